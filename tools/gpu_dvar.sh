# GPU box: decode timing for each COMET_NVCC_DEFS variant given as arguments (commas = spaces).
for defs in "$@"; do
  echo "=== variant: $defs"
  COMET_NVCC_DEFS="${defs//,/ }" timeout 600 python -c "from paper_conf_asplos_liu0rxpwl0w25_b200 import build; build.build(force=True)" > /dev/null 2>&1 || { echo build failed; continue; }
  timeout 300 python tools/decode_time.py --Ms ${DEC_MS:-1,32} --layers ${DEC_LAYERS:-gate_up,qkv} 2>&1 | grep -v "^{"
done
