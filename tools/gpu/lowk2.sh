for c in c5 c3; do for lm in 128 256 512; do MF_UPD_LOWK_MAX=$lm timeout 600 python tools/la_ab.py $c nbranch=4 2>&1 | sed "s/^/lowkmax=$lm /"; done; done
