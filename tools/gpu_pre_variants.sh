# Prefill-kernel compile-time variant sweep on the GPU box (headline GEMM TOPS per variant).
for defs in "$@"; do
  echo "=== variant: [$defs]"
  COMET_NVCC_DEFS="$defs" python -c "from paper_conf_asplos_liu0rxpwl0w25_b200 import build; build.build(force=True)" > /dev/null 2>&1 || { echo build failed; continue; }
  timeout 300 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --cpu-budget 0 --decode 0 --configs 0 ${BENCH_ARGS} 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']
print('achieved', round(r['achieved'],1), 'frac', round(r['frac'],3), {k: round(v) for k,v in r['per_layer_gemm_us'].items()})"
done
