mkdir -p gpurun_out
python scripts/h2d_bw.py > gpurun_out/h2d_bw.txt 2>&1; cat gpurun_out/h2d_bw.txt
