# final build of the session: smoke, default bench line, launch list
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
python bench.py > gpurun_out/r53_bench.json 2> gpurun_out/r53_bench.err; head -c 300 gpurun_out/r53_bench.json; echo
python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/r53_ref.json 2>&1; head -c 200 gpurun_out/r53_ref.json; echo
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r53_launches.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu-baseline --profile-steps 1 > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/r53_launches.csv > gpurun_out/r53_launches_summary.txt 2>&1; tail -15 gpurun_out/r53_launches_summary.txt
