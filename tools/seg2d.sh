# 2D segment-length sweep (wave fill of the C2 grid): MRLBM_SEG for C2 fp64 / fp32
TAG=${1:-seg2d}
mkdir -p gpurun_out
for rep in 1 2; do
for prec in fp64 fp32; do
  for seg in 24 23 22 26 20 32; do
    MRLBM_SEG=$seg timeout 120 python bench.py --config C2 --precision $prec --steps 1000 --no-cpu-baseline --no-e2e \
      | sed "s/^{/{\"lib\": \"seg$seg\", /" >> gpurun_out/${TAG}.jsonl 2>> gpurun_out/${TAG}.err
  done
done
done
python tools/show_ab.py gpurun_out/${TAG}.jsonl
