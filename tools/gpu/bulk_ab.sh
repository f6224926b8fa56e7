set -x
NB=1 timeout 900 python tools/bulk_ab.py c3 0,0r,1,1r,2,3 > gpurun_out/bulk_ab_c3.txt 2>&1; grep mode gpurun_out/bulk_ab_c3.txt
NB=1 timeout 1200 python tools/bulk_ab.py c5 0,1,2,3 > gpurun_out/bulk_ab_c5.txt 2>&1; grep mode gpurun_out/bulk_ab_c5.txt
