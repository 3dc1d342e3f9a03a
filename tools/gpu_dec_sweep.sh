# Decode-kernel compile-time variant sweep (GPU box): builds each variant and times config 5.
for defs in ${VARIANTS:-"" "-DCOMET_DEC_PDL=0" "-DCOMET_WAIT_MODE=2" "-DCOMET_WAIT_MODE=1"}; do
  echo "== variant: [$defs]"
  COMET_NVCC_DEFS="$defs" python -c "from paper_conf_asplos_liu0rxpwl0w25_b200 import build; build.build(force=True)" > /dev/null 2>&1 || { echo build failed; continue; }
  timeout 120 python tools/decode_time.py --Ms 1,8,32 --layers gate_up,qkv --iters 40 2>&1 | tail -7 | head -6
done
