python -c "
import sys; sys.path.insert(0,'.')
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
import torch; torch.cuda.init()
p = torch.cuda.get_device_properties(0)
print('smem/SM', p.shared_memory_per_multiprocessor, 'optin', p.shared_memory_per_block_optin)
for M in (8,32):
  for N,K in ((15360,5120),(5120,5120),(20480,5120),(5120,20480)):
    print(M,N,K,L.gemm_plan(M,N,K))
" > gpurun_out/c3_plans.txt 2>&1
timeout 120 python tools/chain_bench.py 8 >> gpurun_out/c3_chain.txt 2>&1
for S in 2 3 4 5 6 7 8; do LIGER_GEMM_FORCE_SPLITS=$S timeout 120 python tools/chain_bench.py 8 >> gpurun_out/c3_chain.txt 2>&1; done
timeout 300 python tools/pass_timing.py 8 >> gpurun_out/c3_pass.txt 2>&1
