for r in 1 2; do
for b in 8 4; do
 timeout 300 python tools/pass_timing.py $b >> gpurun_out/co_pass.txt 2>&1
 LIGER_NO_CARVEOUT=1 timeout 300 python tools/pass_timing.py $b >> gpurun_out/co_pass_off.txt 2>&1
done; done
