"""CPU oracle for the Liger hot path — TEST INFRASTRUCTURE ONLY.

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s `cpu_baseline` /
`--impl reference` legs may import this package.  The product path
(`paper_conf_ppopp_duwjchcl24_b200`) never imports it and fails loudly when its
CUDA library is missing.  The oracle shares no code with the CUDA path; both
read seeded inputs from `liger_inputs` (generators only, no method arithmetic).

Modules
  model      plain fp64 numpy forward of the (unsharded and TP-sharded)
             decoder layer and the greedy full model
  scheduler  Algorithm 1 with contention factor and runtime decomposition
             (§3.4-3.6)
  metrics    latency / throughput definitions (C11)

Pins (tests/test_oracle_*.py): HF transformers OPTForCausalLM in fp64, closed
forms, brute force on tiny inputs, TP/decomposition/KV-cache invariants, the
hand-worked Algorithm 1 example.  Throughput/latency numbers of the paper are
context only: parity unpinned for them.
"""
