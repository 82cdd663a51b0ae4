set -x
timeout 600 python -m pytest tests/test_gpu_parity.py -k "gemm" -x -q > gpurun_out/c_pytest.log 2>&1; echo rc=$? >> gpurun_out/c_pytest.log
timeout 600 python -m pytest tests/test_gpu_tp_loopback.py -x -q > gpurun_out/c_loop.log 2>&1; echo rc=$? >> gpurun_out/c_loop.log
for M in 2 8 32; do
 timeout 120 python tools/chain_bench.py $M >> gpurun_out/c_chain.txt 2>&1
 LIGER_GEMM_NO_CLUSTER=1 timeout 120 python tools/chain_bench.py $M >> gpurun_out/c_chain_nocl.txt 2>&1
done
python -c "
import sys; sys.path.insert(0,'.')
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
import torch; torch.cuda.init()
for M in (2,8,32):
  for N,K in ((15360,5120),(5120,5120),(20480,5120),(5120,20480)):
    print(M,N,K,L.gemm_plan(M,N,K))
" > gpurun_out/c_plans.txt 2>&1
for b in 2 8; do
 timeout 300 python tools/pass_timing.py $b >> gpurun_out/c_pass.txt 2>&1
 LIGER_GEMM_NO_CLUSTER=1 timeout 300 python tools/pass_timing.py $b >> gpurun_out/c_pass_nocl.txt 2>&1
done
