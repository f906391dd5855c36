# segment-length sweep: 2D (C2 fp64/fp32) shorter segments; 3D (C3, C5w) segment lengths
TAG=${1:-segsweep}
mkdir -p gpurun_out
one() { MRLBM_SEG=$1 timeout 150 python bench.py $2 --steps $3 --no-cpu-baseline --no-e2e | sed "s/^{/{\"lib\": \"seg$1\", /" >> gpurun_out/${TAG}.jsonl 2>> gpurun_out/${TAG}.err; }
for prec in fp64 fp32; do for seg in 20 18 16 14 12 10; do one $seg "--config C2 --precision $prec" 1000; done; done
for seg in 0 24 32 48 64 128; do one $seg "--config C3" 300; done
for seg in 0 16 32 64; do one $seg "--config C5" 100; done
for seg in 0 32 64; do one $seg "--config C4" 100; done
python tools/show_ab.py gpurun_out/${TAG}.jsonl
