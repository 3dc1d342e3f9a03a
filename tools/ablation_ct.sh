# SURVEY §8(d) compile-time ablations of the prefill pair kernel (GPU box): headline GEMM TOPS per
# variant, as JSON lines in $OUT/ablation_ct.jsonl.  Variants: production; B pre-widened by TMA
# (upper bound of skipping the widen work, 2x weight bytes; timing only); scalar FFMA promotion;
# magic-number INT8 conversion; pipeline depth S = 3 (S = 4 is production; 2 and >= 5 do not fit
# the two-accumulator ring / shared memory).
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
: > $OUT/ablation_ct.jsonl
for defs in "" "-DCOMET_PREWIDENED_UB=1" "-DCOMET_PROMO_SCALAR=1" "-DCOMET_I2F_MAGIC=1" "-DCOMET_N256_SMEM_KB=160" ""; do
  COMET_NVCC_DEFS="$defs" python -c "from paper_conf_asplos_liu0rxpwl0w25_b200 import build; build.build(force=True)" > /dev/null 2>&1 || { echo "{\"defs\": \"$defs\", \"error\": \"build failed\"}" >> $OUT/ablation_ct.jsonl; continue; }
  timeout 300 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --cpu-budget 0 --decode 0 --configs 0 2>/dev/null | DEFS="$defs" python -c "
import json, os, sys
d = json.loads(sys.stdin.read().strip().splitlines()[-1]); r = d['roofline']
print(json.dumps({'defs': os.environ['DEFS'], 'gemm_tops': round(r['achieved'], 1), 'frac': round(r['frac'], 4),
                  'us': {k: round(v, 1) for k, v in r['per_layer_gemm_us'].items()}, 'clocks': d['clocks']}))" >> $OUT/ablation_ct.jsonl
done
python -c "from paper_conf_asplos_liu0rxpwl0w25_b200 import build; build.build(force=True)" > /dev/null 2>&1
cat $OUT/ablation_ct.jsonl
