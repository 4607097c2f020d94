#!/bin/bash
# Developer build with the DG_EXP cost-breakdown switches compiled in
# (dg_kernels.cu EXP_ON): paper_conf_asplos_zhangl0hlg19_b200/libdigraph_exp.so,
# loaded with DG_LIB_PATH=<that file>.  Never the product library.
set -e
cd "$(dirname "$0")/.."
DG_NVCC_EXTRA=-DDG_EXP python - <<'PY'
import os
import paper_conf_asplos_zhangl0hlg19_b200.build as b
b.OUT = os.path.join(b.HERE, "libdigraph_exp.so")
b.BUILD = os.path.join(b.HERE, "_build_exp")
print(b.build(force=True))
PY
