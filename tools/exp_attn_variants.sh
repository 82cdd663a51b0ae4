# decode attention ring depth x CTAs per SM variants, each built in a scratch copy of the repo
for v in "4 3" "2 6" "3 4" "2 5"; do
  set -- $v
  d=/tmp/attn_v_$1_$2; rm -rf $d; mkdir -p $d
  cp -r paper_conf_ppopp_duwjchcl24_b200 liger_inputs oracle tools include MEASURED_PEAKS.json $d/ 2>/dev/null
  rm -rf $d/paper_conf_ppopp_duwjchcl24_b200/build $d/paper_conf_ppopp_duwjchcl24_b200/libliger.so
  sed -i "s/constexpr int DC_NS = 4;/constexpr int DC_NS = $1;/; s/constexpr int DC_CTAS_PER_SM = 3;/constexpr int DC_CTAS_PER_SM = $2;/" $d/paper_conf_ppopp_duwjchcl24_b200/csrc/attn_decode.cuh
  (cd $d && python -c "from paper_conf_ppopp_duwjchcl24_b200 import build as b; b.build()" > /dev/null 2>&1) || { echo "build failed $v"; continue; }
  echo "== DC_NS=$1 CTAS_PER_SM=$2"
  (cd $d && timeout 120 python tools/kbench_attn.py 2>&1 | grep attn_decode)
  (cd $d && timeout 200 python tools/pass_timing.py 8 2>&1 | tail -1)
done
