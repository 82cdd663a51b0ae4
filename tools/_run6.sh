for CH in 0 32 64 128; do
 echo "== CH=$CH" >> gpurun_out/a_kb.txt
 LIGER_ATTN_CHUNK=$CH timeout 200 python tools/kbench_attn.py >> gpurun_out/a_kb.txt 2>&1
done
for CH in 0 64 128; do
 for b in 2 8; do
  echo "== CH=$CH" >> gpurun_out/a_pass.txt
  LIGER_ATTN_CHUNK=$CH timeout 300 python tools/pass_timing.py $b >> gpurun_out/a_pass.txt 2>&1
 done
done
