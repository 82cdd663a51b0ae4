timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "fused or fusion or layernorm" > gpurun_out/f_pytest.log 2>&1; echo rc=$? >> gpurun_out/f_pytest.log
for b in 2 8; do
 timeout 300 python tools/pass_timing.py $b >> gpurun_out/f_pass.txt 2>&1
 LIGER_FUSE_SPLITK_LN=0 timeout 300 python tools/pass_timing.py $b >> gpurun_out/f_pass_nofuse.txt 2>&1
done
