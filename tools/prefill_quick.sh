# GPU box: prefill GEMM quick check -- bench headline (no sweeps) + pair-kernel exact tests.
python -c "import __graft_entry__ as g; g.build()" > /dev/null
python bench.py --steps 10 --warmup 3 --e2e-steps 0 --cpu-budget 0 --decode 0 --configs 0 ${BENCH_ARGS} 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']
print('value', round(d['value'],1), 'achieved', round(r['achieved'],1), 'frac', round(r['frac'],3), {k: round(v) for k,v in r['per_layer_gemm_us'].items()})"
timeout 600 python -m pytest tests/test_gpu_exact.py -q -x -k "pair or c4 or c3 or single" 2>&1 | tail -2
