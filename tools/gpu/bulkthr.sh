for c in c5 c4 c3; do
 MF_UPD_BULK_TILES=2368 MF_UPD_BULK_K=512 timeout 600 python tools/la_ab.py $c nbranch=4 2>&1 | sed "s/^/2368,512 /"
 MF_UPD_BULK_TILES=1184 MF_UPD_BULK_K=512 timeout 600 python tools/la_ab.py $c nbranch=4 2>&1 | sed "s/^/1184,512 /"
 MF_UPD_BULK_TILES=2368 MF_UPD_BULK_K=256 timeout 600 python tools/la_ab.py $c nbranch=4 2>&1 | sed "s/^/2368,256 /"
 MF_UPD_BULK_TILES=4736 MF_UPD_BULK_K=1024 timeout 600 python tools/la_ab.py $c nbranch=4 2>&1 | sed "s/^/4736,1024 /"
done
