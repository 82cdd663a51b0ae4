timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/v3_pytest.log 2>&1; echo pytest=$? >> gpurun_out/v3_pytest.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/v3_smoke.log 2>&1
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,temperature.gpu,power.draw --format=csv > gpurun_out/v3_smi.txt
timeout 600 python bench.py > gpurun_out/v3_bench.json 2> gpurun_out/v3_bench.err
timeout 600 python bench.py --workload generative --no-cpu-baseline > gpurun_out/v3_bench_gen.json 2> gpurun_out/v3_bench_gen.err
timeout 600 python bench.py --impl reference > gpurun_out/v3_bench_ref.json 2> gpurun_out/v3_bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -s 700 -c 3000 --csv --log-file gpurun_out/v3_launches_decode_b8.csv python tools/profile_run.py 8 256 4 > gpurun_out/v3_ncu_run.log 2>&1
