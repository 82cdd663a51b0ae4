timeout 900 python -m pytest tests/test_gpu_engine.py tests/test_gpu_tp_loopback.py -q -x > gpurun_out/f2_pytest.log 2>&1; echo rc=$? >> gpurun_out/f2_pytest.log
for b in 2 8; do timeout 300 python tools/pass_timing.py $b >> gpurun_out/f2_pass.txt 2>&1; done
timeout 600 python bench.py --workload generative --no-cpu-baseline --no-latency > gpurun_out/f2_gen.json 2> gpurun_out/f2_gen.err
LIGER_LN_FOLD=0 timeout 600 python bench.py --workload generative --no-cpu-baseline --no-latency > gpurun_out/f2_gen_off.json 2>> gpurun_out/f2_gen.err
