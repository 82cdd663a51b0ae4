timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/v2_pytest.log 2>&1; echo pytest=$? >> gpurun_out/v2_pytest.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/v2_smoke.log 2>&1
timeout 600 python bench.py > gpurun_out/v2_bench.json 2> gpurun_out/v2_bench.err
timeout 600 python bench.py --workload generative --no-cpu-baseline > gpurun_out/v2_bench_gen.json 2> gpurun_out/v2_bench_gen.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/v2_bench_ref.json 2> gpurun_out/v2_bench_ref.err
