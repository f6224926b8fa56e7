for v in 2 4 8 0; do echo "== VAR $v"; MF_UPD_VAR=$v timeout 1500 python tools/bulk_diff.py c3 3 5 2>&1 | grep "^run"; done
