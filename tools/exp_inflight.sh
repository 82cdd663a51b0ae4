set -x
B="python bench.py --no-latency --no-cpu-baseline --quick"
for args in "" "--inflight 3" "--inflight 4"; do
  timeout 300 $B $args > gpurun_out/e1.log 2>&1; python - <<'P' "$args"
import json,sys
l=[x for x in open('gpurun_out/e1.log') if x.startswith('{')]
d=json.loads(l[-1]) if l else {}
print('ARGS',sys.argv[1],d.get('value'),d.get('ms_per_step'),d.get('decode_pass_in_situ',{}).get('us'))
P
done
for r in 8 16; do
  LIGER_GEMM_SM_RESERVE=$r timeout 300 $B > gpurun_out/e1.log 2>&1; python - <<'P' "$r"
import json,sys
l=[x for x in open('gpurun_out/e1.log') if x.startswith('{')]
d=json.loads(l[-1]) if l else {}
print('RSV',sys.argv[1],d.get('value'),d.get('ms_per_step'))
P
done
tail -5 gpurun_out/e1.log
