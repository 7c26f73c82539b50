#!/bin/bash
# existing tuning knobs re-checked against the current defaults (serpentine order changed the memory behaviour)
cd $GRAFT_REPO_ROOT
bash tools/gpu/ab.sh knobs C2 10 2 "-" "panel_tw=32" "panel_pf=0" "trsm=2" "trsm=3" "spmv=17"
bash tools/gpu/ab.sh knobs3 C3 5 1 "-" "panel_tw=32" "panel_pf=0"
