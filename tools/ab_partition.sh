mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gputests16.log 2>&1; tail -1 gpurun_out/gputests16.log
NCU='ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum --clock-control none -k regex:part_ -c 6 --csv'
$NCU --log-file gpurun_out/ab16.csv python tools/profile_run.py --replicas 1024 --seconds 600 --repeat 2 > /dev/null 2>&1
sed -i 's/^constexpr int kSU = 16;/constexpr int kSU = 8; /' paper_conf_middleware_bhasisjgpkd24_b200/csrc/partition.cu
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build8.log 2>&1
$NCU --log-file gpurun_out/ab8.csv python tools/profile_run.py --replicas 1024 --seconds 600 --repeat 2 > /dev/null 2>&1
timeout 300 python bench.py --cpu-sample 0 --e2e-replicas 0 > gpurun_out/bench8.log 2>&1; tail -1 gpurun_out/bench8.log | cut -c1-120
