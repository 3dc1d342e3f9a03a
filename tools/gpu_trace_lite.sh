# Low-overhead pipeline trace of the prefill pair kernel (events 0 producer, 3/11 MMA issue,
# 6 promotion wake, 10 accumulator released, 12 promotion before its wait) on the GPU box:
#   TRACE_DEFS="-D..." bash tools/gpu_trace_lite.sh
COMET_NVCC_DEFS="-DCOMET_TRACE=1 -DCOMET_TRACE_MASK=0x1C49 $TRACE_DEFS" timeout 600 python -c "from paper_conf_asplos_liu0rxpwl0w25_b200 import build; build.build(force=True)" > /dev/null 2>&1
timeout 300 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --cpu-budget 0 --decode 0 --configs 0 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']; print('trace build achieved', round(r['achieved'],1), {k: round(v) for k,v in r['per_layer_gemm_us'].items()})"
timeout 120 python tools/trace_gemm.py 3 > gpurun_out/trace_lite.json && python tools/trace_analyze.py gpurun_out/trace_lite.json 0 2>/dev/null | grep -v "nan"
