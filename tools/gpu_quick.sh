# GPU box: parity tests + decode timing + short bench (GEMM/quantize per layer).
python -c "from paper_conf_asplos_liu0rxpwl0w25_b200 import build; build.build(force=True)" > /dev/null 2>&1
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
timeout 300 python tools/decode_time.py ${DEC_ARGS} 2>&1 | head -14
if [ -z "$NO_BENCH" ]; then
timeout 300 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --cpu-budget 0 --decode 0 2>&1 | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']
print('value', round(d['value'],1), 'achieved', round(r['achieved'],1), 'frac', round(r['frac'],3), {k: round(v,1) for k,v in r['per_layer_gemm_us'].items()}, {k: round(v,1) for k,v in r['per_layer_quantize_us'].items()})"
fi
