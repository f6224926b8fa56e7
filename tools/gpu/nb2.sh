for c in c5 c4 c3 c2; do timeout 600 python tools/la_ab.py $c nbranch=2,4,8 2>&1; done
