mkdir -p gpurun_out/prof2
python __graft_entry__.py > /dev/null 2>&1
ARLO_PROFILE_TIMED=1 timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv \
    --log-file gpurun_out/prof2/launches.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu-baseline \
    > gpurun_out/prof2/bench_under_ncu.log 2>&1
python tools/forward_breakdown.py --summarize gpurun_out/prof2/launches.csv > gpurun_out/prof2/launches_summary.txt 2>&1
timeout 1200 python tools/trace_replay_100k.py 100000 > gpurun_out/prof2/trace_replay_100k.json 2> gpurun_out/prof2/trace_replay_100k.err
