# Round profile artifacts (run on the GPU box from the repo root; OUT defaults to gpurun_out):
#   bench_full.json    default bench.py line (N=1)
#   launches.csv       ncu launch list of a short bench run (cold-cache, serialised)
#   prof_gemm          ncu --set full of the 3 prefill GEMM launches of one step (gate_up, down, qkv)
#   prof_quant         ncu --set full of the 3 quantize launches of one step
#   prof_dec / prof_fixup  TMEM decode GEMM (orientation 1, LLaMA-3-70B gate/up, M=1) and its fix-up kernel
#   prof_gemv          warp-level decode GEMM (orientation 4, the auto plan there) and its reduction kernel
#   prof_perm / prof_kv4   NEXT-1 fused-permutation quantise, NEXT-4 KV4 kernels
OUT=${OUT:-gpurun_out}
set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 900 python bench.py > $OUT/bench_full.json 2> $OUT/bench_full.err; tail -c 2000 $OUT/bench_full.json
SHORT="python bench.py --steps 2 --warmup 3 --e2e-steps 0 --cpu-budget 0 --decode 0 --configs 0"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $OUT/launches.csv $SHORT > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_w4ax_n -s 3 -c 3 -f -o $OUT/prof_gemm $SHORT > $OUT/prof_gemm.log 2>&1; tail -2 $OUT/prof_gemm.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_quantize -s 6 -c 3 -f -o $OUT/prof_quant $SHORT > $OUT/prof_quant.log 2>&1; tail -2 $OUT/prof_quant.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:^k_w4ax$ -s 2 -c 1 -f -o $OUT/prof_dec python tools/decode_time.py --Ms 1 --layers gate_up --iters 2 --orientation 1 > $OUT/prof_dec.log 2>&1; tail -2 $OUT/prof_dec.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_fixup -s 2 -c 1 -f -o $OUT/prof_fixup python tools/decode_time.py --Ms 1 --layers gate_up --iters 2 --orientation 1 > $OUT/prof_fixup.log 2>&1; tail -2 $OUT/prof_fixup.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_gemv -s 4 -c 2 -f -o $OUT/prof_gemv python tools/decode_time.py --Ms 1 --layers gate_up --iters 2 --orientation 4 > $OUT/prof_gemv.log 2>&1; tail -2 $OUT/prof_gemv.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_quantize_perm -s 1 -c 1 -f -o $OUT/prof_perm python tools/perm_prof.py 8192 > $OUT/prof_perm.log 2>&1; tail -1 $OUT/prof_perm.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_kv4 -s 2 -c 2 -f -o $OUT/prof_kv4 python tools/kv4_prof.py > $OUT/prof_kv4.log 2>&1; tail -1 $OUT/prof_kv4.log
for r in gemm quant dec fixup gemv perm kv4; do python tools/ncu_summary.py $OUT/prof_$r.ncu-rep > $OUT/ncu_${r}_full.json 2>/dev/null; done
ls -la $OUT
