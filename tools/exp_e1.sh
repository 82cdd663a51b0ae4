# E1 placement: loopback TP = 2 bench dry run (functional; timing shared by two ranks on one GPU)
for lead in -1 0 20 60; do
  LIGER_E1_LEAD_US=$lead timeout 600 python bench.py --gpus 2 --loopback --quick --no-latency --steps 4 --warmup 3 > gpurun_out/e1.log 2>&1
  python - "$lead" <<'P'
import json,sys
l=[x for x in open('gpurun_out/e1.log') if x.startswith('{')]
d=json.loads(l[-1]) if l else {}
print('LEAD', repr(sys.argv[1]), d.get('value'), d.get('host'))
P
done
timeout 600 python -m pytest tests/test_gpu_tp_loopback.py -x -q 2>&1 | tail -2
