# round-2 measurement session: bench lines for every config (MR + ST), side runs, reference arm, ncu
TAG=${1:-r02b}
mkdir -p gpurun_out
timeout 300 python tools/p2p_overhead.py > gpurun_out/${TAG}_p2p_overhead.json 2> gpurun_out/${TAG}_p2p_overhead.err; cat gpurun_out/${TAG}_p2p_overhead.json
timeout 900 python bench.py > gpurun_out/${TAG}_default.json 2> gpurun_out/${TAG}_default.err; tail -c 300 gpurun_out/${TAG}_default.err
for cfg in "C2 fp32" "C3 fp64" "C4 fp32" "C5 fp64"; do set -- $cfg
  timeout 400 python bench.py --config $1 --precision $2 >> gpurun_out/${TAG}_all.jsonl 2>> gpurun_out/${TAG}_all.err
done
for cfg in "C2 fp64" "C3 fp64" "C4 fp32"; do set -- $cfg
  timeout 400 python bench.py --config $1 --precision $2 --method ST --no-cpu-baseline >> gpurun_out/${TAG}_st.jsonl 2>> gpurun_out/${TAG}_st.err
done
MRLBM_TILE=2 timeout 300 python bench.py --config C5 --steps 200 --no-cpu-baseline | sed 's/^{/{"lib": "tile2_32x16", /' >> gpurun_out/${TAG}_side.jsonl 2>> gpurun_out/${TAG}_side.err
timeout 900 python bench.py --config C5 --strong --steps 40 --warmup 4 --no-cpu-baseline --no-e2e | sed 's/^{/{"lib": "C5_1024cubed_1gpu", /' >> gpurun_out/${TAG}_side.jsonl 2>> gpurun_out/${TAG}_side.err
timeout 600 python bench.py --impl reference --steps 20 --warmup 3 > gpurun_out/${TAG}_reference.json 2> gpurun_out/${TAG}_reference.err
python tools/show_bench.py gpurun_out/${TAG}_default.json gpurun_out/${TAG}_all.jsonl gpurun_out/${TAG}_st.jsonl gpurun_out/${TAG}_side.jsonl
NO_LAUNCHES= bash tools/ncu_capture.sh ${TAG} "C2 fp64" "C2 fp32" "C3 fp64" "C4 fp32" "C5 fp64" > /dev/null 2>&1
ls gpurun_out | grep ${TAG} | head -50
