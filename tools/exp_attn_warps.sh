# decode attention compute warps x CTAs per SM (x ring stages), each built in a scratch copy
for v in "128 3 4" "256 2 4" "192 3 4" "256 2 3"; do
  set -- $v
  d=/tmp/attn_w_$1_$2_$3; rm -rf $d; mkdir -p $d
  cp -r paper_conf_ppopp_duwjchcl24_b200 liger_inputs oracle tools include MEASURED_PEAKS.json $d/ 2>/dev/null
  rm -rf $d/paper_conf_ppopp_duwjchcl24_b200/build $d/paper_conf_ppopp_duwjchcl24_b200/libliger.so
  sed -i "s/constexpr int DC_THREADS = 128;/constexpr int DC_THREADS = $1;/; s/constexpr int DC_CTAS_PER_SM = 3;/constexpr int DC_CTAS_PER_SM = $2;/; s/constexpr int DC_NS = 4;/constexpr int DC_NS = $3;/" $d/paper_conf_ppopp_duwjchcl24_b200/csrc/attn_decode.cuh
  (cd $d && python -c "from paper_conf_ppopp_duwjchcl24_b200 import build as b; b.build()" > /dev/null 2>&1) || { echo "build failed $v"; continue; }
  echo "== threads=$1 ctas/SM=$2 stages=$3 $(cuobjdump --dump-resource-usage $d/paper_conf_ppopp_duwjchcl24_b200/libliger.so 2>/dev/null | grep -A1 'attn_decode_kernelILi128' | grep -o 'REG:[0-9]* STACK:[0-9]*')"
  (cd $d && timeout 120 python tools/kbench_attn.py 2>&1 | grep attn_decode)
  (cd $d && timeout 200 python tools/pass_timing.py 8 2>&1 | tail -1)
done
