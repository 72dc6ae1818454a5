mkdir -p gpurun_out
for lc in 0 74 100 128; do
 timeout 300 python scripts/sweep.py --opt leaf_ctas=$lc --opt leaf_width=32,48,64 >> gpurun_out/sweep.log 2>&1 || echo "fail lc=$lc" >> gpurun_out/sweep.log
done
timeout 300 python scripts/leaf_scan.py >> gpurun_out/sweep.log 2>&1
cat gpurun_out/sweep.log | grep -v Warn
