O=gpurun_out/p3; mkdir -p $O
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_eval3w -c 1 -o $O/k3w_k1 python tools/profile3d.py 8000 1 > $O/ncu.log 2>&1
python tools/ncu_summary.py $O/k3w_k1.ncu-rep > $O/summary.txt 2>&1
head -120 $O/summary.txt
