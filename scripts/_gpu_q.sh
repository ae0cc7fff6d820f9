mkdir -p gpurun_out/q
OUT=gpurun_out/q STEPS=20 SPECS="--config cd" KNOBS="|--gring 10 --variant 9|--gring 10|--gring 10 --variant 9 --branches 3" bash scripts/knob_sweep.sh > /dev/null 2>&1
cat gpurun_out/q/sweep.log
