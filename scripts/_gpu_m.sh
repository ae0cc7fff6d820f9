mkdir -p gpurun_out/m
OUT=gpurun_out/m STEPS=20 SPECS="--config c5|--config c3" KNOBS="|--variant 7|--variant 8" bash scripts/knob_sweep.sh > /dev/null 2>&1
cat gpurun_out/m/sweep.log
