#!/bin/bash
# dev: run the determinism probe against the SPMV_DEBUG_WINDOW build
cd paper_conf_ispass_balajicjk23_b200 && cp libspmv.so /tmp/libspmv_rel.so && cp libspmv_dbg.so libspmv.so && cd ..
python scripts/debug_determinism.py 2>&1 | head -40
