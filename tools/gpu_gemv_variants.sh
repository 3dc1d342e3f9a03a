# orientation-4 decode kernel (gemm_v.cu) compile-time variant sweep on the GPU box
for defs in "$@"; do
  echo "=== variant: [$defs]"
  COMET_NVCC_DEFS="$defs" python -c "from paper_conf_asplos_liu0rxpwl0w25_b200 import build; build.build(force=True)" > /dev/null 2>&1 || { echo build failed; continue; }
  timeout 300 python tools/gemv_ab.py ${ORIENTS:-4}
done
