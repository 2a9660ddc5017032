mkdir -p gpurun_out
( AP_EXP_FRAMES=4096,64,65,66,72,80,96,64 AP_EXP_GRIDS=64,148 timeout 600 python tools/exp_c1.py ) > gpurun_out/r2_exp_c1b.txt 2>&1
