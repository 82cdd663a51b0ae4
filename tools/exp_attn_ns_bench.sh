# decode attention ring depth in the two-stream capacity run: scratch builds, bench.py --quick capacity
for ns in 4 3; do
  d=/tmp/attn_ns_$ns; rm -rf $d; mkdir -p $d
  cp -r paper_conf_ppopp_duwjchcl24_b200 liger_inputs oracle tools include bench.py MEASURED_PEAKS.json profiles $d/ 2>/dev/null
  rm -rf $d/paper_conf_ppopp_duwjchcl24_b200/build $d/paper_conf_ppopp_duwjchcl24_b200/libliger.so
  sed -i "s/constexpr int DC_NS = 4;/constexpr int DC_NS = $ns;/" $d/paper_conf_ppopp_duwjchcl24_b200/csrc/attn_decode.cuh
  (cd $d && python -c "from paper_conf_ppopp_duwjchcl24_b200 import build as b; b.build(); b.build_oracle()" > /dev/null 2>&1) || echo "build failed $ns"
done
for i in 1 2; do for ns in 4 3; do
  (cd /tmp/attn_ns_$ns && timeout 300 python bench.py --no-latency --no-cpu-baseline --quick > /tmp/ns_$ns.log 2>&1)
  python - $ns <<'P'
import json,sys
l=[x for x in open(f'/tmp/ns_{sys.argv[1]}.log') if x.startswith('{')]
d=json.loads(l[-1]) if l else {}
print('RUN DC_NS', sys.argv[1], d.get('value'), d.get('e2e',{}).get('value'), d.get('decode_pass_in_situ',{}).get('us'))
P
done; done
