# Round profile artifacts (run on the GPU box from the repo root):
#   gpurun_out/bench_full.json   default bench.py line (N=1)
#   gpurun_out/launches.csv      ncu launch list of a short bench run (cold-cache, serialised)
#   gpurun_out/prof_gemm.ncu-rep ncu --set full of the 3 GEMM launches of one step (gate_up, down, qkv)
#   gpurun_out/prof_quant.ncu-rep ncu --set full of the 3 quantize launches of one step
set -x
timeout 600 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; tail -c 3000 gpurun_out/bench_full.json
SHORT="python bench.py --steps 2 --warmup 3 --e2e-steps 0 --cpu-budget 0 --decode 0"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches.csv $SHORT > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_w4ax -s 3 -c 3 -f -o gpurun_out/prof_gemm $SHORT > gpurun_out/prof_gemm.log 2>&1; tail -2 gpurun_out/prof_gemm.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_quantize -s 6 -c 3 -f -o gpurun_out/prof_quant $SHORT > gpurun_out/prof_quant.log 2>&1; tail -2 gpurun_out/prof_quant.log
# decode GEMM (LLaMA-3-70B gate/up, M=1): one ncu --set full capture
timeout 600 ncu --set full --clock-control none --import-source on -k regex:^k_w4ax$ -s 2 -c 1 -f -o gpurun_out/prof_dec python tools/decode_time.py --Ms 1 --layers gate_up --iters 2 > gpurun_out/prof_dec.log 2>&1; tail -2 gpurun_out/prof_dec.log
# NEXT rows: fused-permutation quantise (K = 8192, M = 4096) and the two KV4 kernels
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_quantize_perm -s 1 -c 1 -f -o gpurun_out/prof_perm python tools/perm_prof.py 8192 > gpurun_out/prof_perm.log 2>&1; tail -1 gpurun_out/prof_perm.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_kv4 -s 2 -c 2 -f -o gpurun_out/prof_kv4 python tools/kv4_prof.py > gpurun_out/prof_kv4.log 2>&1; tail -1 gpurun_out/prof_kv4.log
