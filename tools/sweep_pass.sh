#!/bin/bash
# Dev: decode-pass time (tools/pass_timing.py) over environment settings; one line each.
#   bash tools/sweep_pass.sh "B_LIST" "ENV1" "ENV2" ...   (ENV = "" for the defaults, or "K=V K2=V2")
bs="$1"; shift
for cfg in "$@"; do
  for b in $bs; do
    env $cfg timeout 300 python tools/pass_timing.py $b 2>&1 | tail -1 | sed "s/^/[$cfg] /"
  done
done
