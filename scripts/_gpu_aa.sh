mkdir -p gpurun_out/aa
OUT=gpurun_out/aa STEPS=20 SPECS="--config cd" KNOBS="|--gring 10 --variant 9|--gring 10 --variant 5" bash scripts/knob_sweep.sh > /dev/null 2>&1
cat gpurun_out/aa/sweep.log
