# round 2, call b: GPU tests after the saint reservation / low-memory / emulated-rank changes,
# GraphSAINT spike check (6 runs), L2 eviction-hint microbenchmark, papers100M one-rank emulation
set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r2b_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2b_pytest.txt
for i in 1 2 3 4 5 6; do timeout 300 python bench.py --saint --steps 20 --warmup 5 --no-cpu-baseline >> gpurun_out/r2b_saint.jsonl 2>> gpurun_out/r2b_saint.err; done
timeout 600 tools/gather_hint_bench > gpurun_out/r2b_hint.jsonl 2> gpurun_out/r2b_hint.err
timeout 1800 python bench.py --emulate 8 --steps 5 --warmup 3 > gpurun_out/r2b_papers_emul.json 2> gpurun_out/r2b_papers_emul.err
echo done
