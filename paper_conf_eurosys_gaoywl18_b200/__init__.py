"""B200-native cellular batching (BatchMaker, EuroSys'18): the C-ABI library libbm.so
(include/bm.h: C++ scheduler + sm_100a kernels) and its thin Python binding
`paper_conf_eurosys_gaoywl18_b200.bm` (importing it raises if libbm.so is missing: there is
no fallback). `paper_conf_eurosys_gaoywl18_b200.build` compiles the library."""
