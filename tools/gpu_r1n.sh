mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_dist.py -x -q 2>&1 | tail -15
for lr in 0.1 1.0 10.0; do
timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 --ttp-megabatches 40 --lr-max $lr 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); t=d['time_to_p1']; print('lr', t['lr_max'], 'ttp', t['value'], 'best', t['p1_best'], 'floor', t['p1_floor'], t['curve_every_4'])"
done
