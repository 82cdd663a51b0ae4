B="python bench.py --no-latency --no-cpu-baseline --quick"
run() { tag=$1; shift; env "$@" timeout 300 $B > gpurun_out/e2.log 2>&1; python - "$tag" <<'P'
import json,sys
l=[x for x in open('gpurun_out/e2.log') if x.startswith('{')]
d=json.loads(l[-1]) if l else {}
print('RUN',sys.argv[1],d.get('value'),d.get('ms_per_step'),d.get('decode_pass_in_situ',{}).get('us'))
P
}
run base X=1
run nopdl LIGER_NO_PDL=1
run serial_streams LIGER_T1_STREAMS=0
run serial_nopdl LIGER_T1_STREAMS=0 LIGER_NO_PDL=1
LIGER_NO_PDL=1 timeout 400 python tools/timeline_capacity.py 4 interleaved 2>&1 | tail -9
