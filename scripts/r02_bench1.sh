#!/bin/bash
O=gpurun_out/r02y; mkdir -p $O
( time timeout 900 python bench.py > $O/bench_c2.log 2>&1 ) 2> $O/time_c2.txt
timeout 600 python bench.py --config c1 --no-e2e > $O/bench_c1.log 2>&1
timeout 600 python bench.py --config c4 > $O/bench_c4.log 2>&1
timeout 600 python bench.py --config c3 --no-sweep > $O/bench_c3.log 2>&1
timeout 600 python bench.py --config c5 > $O/bench_c5.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $O/ref_c2.log 2>&1
tail -c 3000 $O/bench_c2.log; cat $O/time_c2.txt
