for c in c2 c3; do timeout 600 python tools/la_ab.py $c nbranch=2,4,6,8,12; done
