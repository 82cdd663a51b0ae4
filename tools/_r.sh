timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/v5_pytest.log 2>&1; echo pytest=$? >> gpurun_out/v5_pytest.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/v5_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/v5_bench.json 2> gpurun_out/v5_bench.err
timeout 600 python bench.py --workload generative --no-cpu-baseline > gpurun_out/v5_bench_gen.json 2> gpurun_out/v5_bench_gen.err
