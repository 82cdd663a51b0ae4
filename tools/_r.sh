LIGER_T1_STREAMS=1 timeout 900 python bench.py --no-cpu-baseline --no-latency > gpurun_out/t2_on.json 2> gpurun_out/t2.err
timeout 900 python bench.py --no-cpu-baseline --no-latency > gpurun_out/t2_off.json 2>> gpurun_out/t2.err
LIGER_T1_STREAMS=1 LIGER_GEMM_SM_RESERVE=40 timeout 900 python bench.py --no-cpu-baseline --no-latency > gpurun_out/t2_on_r40.json 2>> gpurun_out/t2.err
LIGER_T1_STREAMS=1 LIGER_GEMM_SM_RESERVE=74 timeout 900 python bench.py --no-cpu-baseline --no-latency > gpurun_out/t2_on_r74.json 2>> gpurun_out/t2.err
