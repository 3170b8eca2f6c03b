"""CPU ORACLE for the DGCL halo-exchange hot path — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may import
anything under oracle/.  The product path (paper_conf_eurosys_cai0wmcy21_b200) never imports it and
has no CPU fallback.  The oracle shares no code with the C++/CUDA library: it consumes only the
seeded inputs produced by synth/ (graph, partition, required lists, hash-defined values, topology
descriptors).

Modules (each function cites the PAPER.md passage it follows; "P:n" = /root/reference/PAPER.md
line n):
  halo.py        re-indexing (§4.1), forward graphAllgather (§4.2), backward flat and tree order
                 (§6.1, §6.2), brute-force required sets (§4.1)
  cost.py        the staged cost model t(S) (§5.1 rules)
  spst.py        reference SPST (Algorithm 1) with incrementalLinkCost (Algorithm 2), §5.2
  invariants.py  plan invariants (trees, exactly-once delivery, links exist, cost recomputation)

Pins (tests/test_oracle_*.py, -m "not gpu"): literal worked examples (tests/golden/), closed forms
(G=1, L=0 => out[u] = |D_u|), integer-valued exactness, the complete-relation special case against
torch.distributed all_gather / all_reduce, brute force on tiny graphs, the Fig. 6 planner example.
Parity status of SPST beyond the worked example: partially pinned (exact plans are pinned only by
the worked example and derived properties).
"""
