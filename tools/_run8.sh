timeout 600 python -m pytest tests/test_gpu_tp_loopback.py -q -x > gpurun_out/sm_pytest.log 2>&1; echo rc=$? >> gpurun_out/sm_pytest.log
timeout 900 python bench.py --steps 6 --warmup 3 --no-latency --no-cpu-baseline > gpurun_out/sm_bench.json 2> gpurun_out/sm_bench.err
