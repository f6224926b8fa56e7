for c in c2 c3 c4 c5; do timeout 600 python tools/la_ab.py $c model=0,1 nbranch=4 2>&1; done
