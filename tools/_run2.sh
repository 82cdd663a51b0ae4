python -c "
import sys; sys.path.insert(0,'.')
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
import torch; torch.cuda.init()
for M in (2,8,32,64):
  for N,K in ((15360,5120),(5120,5120),(20480,5120),(5120,20480),(3456,9216),(9216,1152),(4608,9216),(9216,4608)):
    print(M,N,K,L.gemm_plan(M,N,K))
" > gpurun_out/c2_plans.txt 2>&1
for M in 2 8 32; do
 timeout 120 python tools/chain_bench.py $M >> gpurun_out/c2_chain.txt 2>&1
done
for S in 2 3 4 5 6 7 8; do LIGER_GEMM_FORCE_SPLITS=$S timeout 120 python tools/chain_bench.py 8 >> gpurun_out/c2_chain_forced.txt 2>&1; done
for b in 2 8; do
 timeout 300 python tools/pass_timing.py $b >> gpurun_out/c2_pass.txt 2>&1
done
timeout 600 python -m pytest tests/test_gpu_parity.py -k "gemm" -x -q > gpurun_out/c2_pytest.log 2>&1; echo rc=$? >> gpurun_out/c2_pytest.log
