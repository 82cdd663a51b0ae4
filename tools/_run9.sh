timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/v4_pytest.log 2>&1; echo pytest=$? >> gpurun_out/v4_pytest.log
for b in 2 8; do timeout 300 python tools/pass_timing.py $b >> gpurun_out/v4_pass.txt 2>&1; done
timeout 200 python tools/kbench_attn.py > gpurun_out/v4_kbattn.txt 2>&1
timeout 900 python bench.py > gpurun_out/v4_bench.json 2> gpurun_out/v4_bench.err
