run() { tag=$1; shift; timeout 300 python bench.py --no-latency --no-cpu-baseline --quick "$@" > gpurun_out/e3.log 2>&1; python - "$tag" <<'P'
import json,sys
l=[x for x in open('gpurun_out/e3.log') if x.startswith('{')]
d=json.loads(l[-1]) if l else {}
print('RUN',sys.argv[1],d.get('value'),d.get('e2e',{}).get('value'),d.get('ms_per_step'),d.get('decode_pass_in_situ',{}).get('us'), d.get('host'))
P
}
run base
run inflight3 --inflight 3
timeout 400 python tools/timeline_capacity.py 4 interleaved 2>&1 | tail -10
timeout 600 python -m pytest tests/test_gpu_engine.py -x -q 2>&1 | tail -3
