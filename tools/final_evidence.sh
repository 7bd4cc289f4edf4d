# The round's final on-box evidence (run under gpurun from the repo root): smoke, the
# hash-stamped ncu traffic of the dominant kernels, the bench line and the reference arm,
# the ncu launch list of the bench command, the paper sweeps, and the GPU test suite.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/f_smi.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('SMOKE OK')" > gpurun_out/f_smoke.txt 2>&1
timeout 900 python tools/ncu_traffic.py > gpurun_out/f_ncu_traffic.log 2>&1
python bench.py > gpurun_out/f_bench.json 2> gpurun_out/f_bench.err
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/f_bench_ref.json 2> gpurun_out/f_bench_ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/f_launches_full600.csv python bench.py --steps 2 --warmup 3 > gpurun_out/f_ncu_bench.log 2>&1
timeout 300 python tools/paper_sweep.py g1 10 30 > gpurun_out/f_sweep_g1.jsonl 2>&1
timeout 300 python tools/paper_sweep.py batch 10 > gpurun_out/f_sweep_batch.jsonl 2>&1
[ "$1" = "tests" ] && python -m pytest tests -m gpu -q > gpurun_out/f_gputests.txt 2>&1
tail -2 gpurun_out/f_smoke.txt; tail -3 gpurun_out/f_ncu_traffic.log; tail -2 gpurun_out/f_gputests.txt 2>/dev/null
