# Time bench.py's GEMMs for each "tile_w[:orientation]" given.
for spec in "$@"; do
  tw=${spec%%:*}; orient=0; [ "$spec" != "$tw" ] && orient=${spec#*:}
  timeout 300 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --cpu-budget 0 --tile-w $tw --orientation $orient 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']
print('tile_w $tw orientation $orient', round(r['achieved'],1), round(r['frac'],3), {k: round(v) for k,v in r['per_layer_gemm_us'].items()})"
done
