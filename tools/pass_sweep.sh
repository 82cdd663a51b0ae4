#!/bin/bash
# dev: decode-pass time and the marginal cost of each op class (LIGER_DBG_SKIP; wrong results)
for b in 2 4 8; do python tools/pass_timing.py $b 2>/dev/null; done
for sk in attn ln1,ln2 out qkv fc1 fc2 ln1,ln2,attn; do
  echo -n "skip=$sk: "; LIGER_DBG_SKIP=$sk python tools/pass_timing.py 8 2>/dev/null
done
