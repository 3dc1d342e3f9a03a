# GPU-box check: parity tests, a short bench, and (optional) a diagnostic pipeline trace.
set -x
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 300 python bench.py --steps 20 --warmup 5 --e2e-steps 2 --cpu-budget 2 > gpurun_out/bench_last.json 2> gpurun_out/bench_last.err; tail -c 1200 gpurun_out/bench_last.json; tail -3 gpurun_out/bench_last.err
if [ -n "$TRACE" ]; then
  COMET_NVCC_DEFS="-DCOMET_TRACE=1 $TRACE_DEFS" timeout 600 python -c "from paper_conf_asplos_liu0rxpwl0w25_b200 import build; build.build(force=True)" > /dev/null 2>&1
  timeout 300 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --cpu-budget 0 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('trace build achieved', round(d['roofline']['achieved'],1))"
  timeout 120 python tools/trace_gemm.py 3 > gpurun_out/trace_last.json && python tools/trace_analyze.py gpurun_out/trace_last.json 0
fi
if [ -n "$PROF" ]; then
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_w4ax_n -c 1 -o gpurun_out/prof_cur -f python bench.py --steps 1 --warmup 0 --e2e-steps 0 --cpu-budget 0 > gpurun_out/prof_cur.log 2>&1; tail -2 gpurun_out/prof_cur.log
fi
