#!/bin/bash
# Round-2 GPU session B: feed-pipeline probe, timeline, Crush-scale battery,
# feed scaling, fill A/B, ncu launch list + full capture (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python tools/lr_feed_probe.py "" "GG_FEED_CHUNK_MB=8" "GG_FEED_CHUNK_MB=32" "GG_FEED_CHUNKS=8" \
  "HOST_THREADS=12" "HOST_THREADS=8" "GG_FEED_NO_NT=1" > gpurun_out/lr_feed_probe.json 2> gpurun_out/lr_feed_probe.err
timeout 600 python tools/timeline.py > gpurun_out/timeline.json 2> gpurun_out/timeline.err
timeout 900 python tools/feed_scaling.py --ranks 1 2 4 8 --same-gpu > gpurun_out/feed_scaling.json 2> gpurun_out/feed_scaling.err
AB_REPS=3 timeout 900 python tools/ab_fill.py "" "GG_FILL_PAIR=1" "GG_FILL_PAIR=3" "GG_FILL_PAIR=4" > gpurun_out/ab_fill.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-ondemand --no-apps > gpurun_out/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gg_fill64 -s 1 -c 1 \
  -o gpurun_out/prof_fill python tools/prof_fill.py > gpurun_out/ncu_full.log 2>&1
timeout 2400 python tools/battery_big.py > gpurun_out/battery.json 2> gpurun_out/battery.err
exit 0
