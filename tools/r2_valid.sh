# round-2 validation: full GPU suite, smoke, sanitizers, P2P overhead
TAG=${1:-r02v}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.max.sm,power.limit --format=csv > gpurun_out/${TAG}_smi.txt 2>&1
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1 || { echo "smoke failed"; tail -5 gpurun_out/${TAG}_smoke.log; exit 1; }
timeout 1500 python -m pytest tests -q -m gpu --timeout 300 > gpurun_out/${TAG}_pytest.log 2>&1; tail -3 gpurun_out/${TAG}_pytest.log
timeout 300 python tools/p2p_overhead.py > gpurun_out/${TAG}_p2p_overhead.json 2> gpurun_out/${TAG}_p2p_overhead.err; cat gpurun_out/${TAG}_p2p_overhead.json
bash tools/sanitize.sh 2>&1 | tee gpurun_out/${TAG}_sanitize_summary.txt
