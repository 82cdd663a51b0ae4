# bench.py --quick capacity runs under experiment knobs (env VAR=value ... per line)
run() { tag=$1; shift; env "$@" timeout 300 python bench.py --no-latency --no-cpu-baseline --quick --workload generative > gpurun_out/ek.log 2>&1; python - "$tag" <<'P'
import json,sys
l=[x for x in open('gpurun_out/ek.log') if x.startswith('{')]
d=json.loads(l[-1]) if l else {}
print('RUN',sys.argv[1],d.get('value'),d.get('e2e',{}).get('value'),d.get('ms_per_step'),d.get('decode_pass_in_situ',{}).get('us'))
P
}
while read -r line; do [ -n "$line" ] && run "$line" $line; done < "${1:-/dev/stdin}"
