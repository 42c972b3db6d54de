"""fp64 CPU oracle for cellular batching (BatchMaker, EuroSys'18).

TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline
and --impl reference legs may import anything under oracle/. The product path (include/bm.h,
the libbm.so C-ABI library and its Python binding in paper_conf_eurosys_gaoywl18_b200/)
never imports, calls or links it, and the oracle shares no code with it: only the seeded
input generators in workloads/ serve both.

  oracle.cells      - one request alone, step by step, float64 (LSTM, Seq2Seq, TreeLSTM)
  oracle.batched    - fp64 batched executor used to brute-force batching equivalence (P4)
  oracle.scheduler  - Algorithm 1 + request processor + slot pool replay in virtual time
"""
