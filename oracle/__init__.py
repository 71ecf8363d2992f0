"""ORACLE — test infrastructure only.

A plain, slow, obviously-correct CPU implementation of what the Mario hot path computes
(PAPER.md: Mario, PPoPP'25). Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s
`cpu_baseline` / `--impl reference` legs may import or execute anything in this package.
The product (`paper_conf_ppopp_liultj25_b200/`, `libmario.so`) never imports it and shares
no code with it; the only shared module is `synth` (seeded inputs, no method arithmetic).

Modules
- `oracle.model`    — decoder LM loss + per-parameter gradients, unpipelined, no
                       checkpointing. Mario reaches exactly this result
                       because checkpointing only replays the forward and the
                       pipeline is synchronous.
- `oracle.schedule` — independent pipeline-schedule oracle: base schedules, the four graph
                       passes, the virtual-pipeline dependency rules (Alg. 1,
                       P:232-240) and the dynamic-programming timeline and
                       memory simulation, written step by step in the paper's order.
- `oracle.replay`   — executes a plan's per-device instruction lists on the CPU with
                       FW/CFW/RC/BW semantics (pins pipelining semantics).

Pins (tests/test_oracle_*.py, tests/test_schedule_oracle.py): central finite differences in
fp64, a torch-fp64 autograd cross-check, closed-form special cases, invariants, and the
paper's Fig. 2 totals (21t/28t/25t/23t/22t). See DESIGN.md "Oracle pins".
"""
