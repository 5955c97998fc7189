#!/bin/bash
# Every round-2 measurement of the current tree on one B200 (run through gpurun):
#   /usr/local/graft/bin/gpurun --timeout 3000 -- 'bash tools/gpu_final.sh'
# Outputs land in gpurun_out/final/; tools/traffic_json.py and tools/ncu_summary.py
# turn them into the committed profiles/ files.
set -x
O=gpurun_out/final
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > $O/smi.txt
python -c "import bench; print(bench._lib_sha())" > $O/sass_sha.txt
timeout 900 python -m pytest tests -m gpu -x -q > $O/gputests.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
# ncu captures of the same library (traffic + stall summary), then the bench (which reads the traffic file)
ncu --set full --clock-control none --import-source on -k regex:k_persistent -s 1 -c 1 -f -o $O/prof_C4 \
    python tools/prof_one.py C4 > $O/ncu_full.log 2>&1
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_atom.sum,lts__t_sectors_srcunit_tex_op_red.sum \
    --clock-control none -k regex:k_persistent -s 1 -c 1 --csv --log-file $O/ncu_window_off.csv \
    python tools/prof_one.py C4 l2_persist=0 > $O/ncu_off.log 2>&1
python tools/traffic_json.py $O > $O/traffic.log 2>&1 && cp profiles/ncu_traffic_C4.json $O/ 
python bench.py > $O/bench.json 2> $O/bench.err
python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-mpm --no-configs > $O/launches.log 2>&1
python tools/cta_trace.py fin C1 C2 C3 C4 > $O/trace.log 2>&1
python tools/phase_breakdown.py fin C1 C2 C3 C4 > $O/phase_breakdown.json 2> $O/phase_breakdown.err
if [ -n "$FULL" ]; then
  # the paper's Table II variants (build them first: bash tools/build_variants.sh tools/variants_f4.txt)
  python tools/ablation_r2.py > $O/ablation_r2.json 2> $O/ablation.err
  python tools/c5_run.py > $O/c5.log 2>&1; cp gpurun_out/c5.json $O/c5_r2.json 2>/dev/null
fi
