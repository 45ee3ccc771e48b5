cd "$(dirname "$0")/.."
python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py > /dev/null 2>&1
timeout 300 python -m pytest tests/test_gpu_round2.py -x -q -m gpu -k "fused_stem or halo" 2>&1 | tail -2
for b in 4 8; do
  timeout 900 python bench.py --bits $b --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --tune --save-plans plans/resnet50_trunk_a${b}_b256.json --layers-json gpurun_out/tune_layers_a$b.json > gpurun_out/tune_a$b.json 2> gpurun_out/tune_a$b.err
  python -c "import json;d=json.load(open('gpurun_out/tune_a$b.json'));print('trunk tuned', $b, d['ms_per_step'], d['parity']['bit_exact'], {k:round(v['us']) for k,v in d['roofline']['families'].items()})"
  cp plans/resnet50_trunk_a${b}_b256.json gpurun_out/tune_plans_a$b.json
done
