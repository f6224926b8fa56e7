for c in c5 c3 c4; do for m in 0 1 2; do MF_UPD_MID=$m timeout 600 python tools/la_ab.py $c nbranch=4 2>&1 | sed "s/^/mid=$m /"; done; done
