# Kernel-1 compile-time variants on the GPU box: tools/quant_bench.py per variant.
for defs in "$@"; do
  echo "=== variant: [$defs]"
  COMET_NVCC_DEFS="$defs" python -c "from paper_conf_asplos_liu0rxpwl0w25_b200 import build; build.build(force=True)" > /dev/null 2>&1 || { echo build failed; continue; }
  timeout 300 python tools/quant_bench.py > /tmp/qb.txt 2>&1; head -2 /tmp/qb.txt
done
