for p in fp32 bf16; do
  for i in 1 2; do timeout 600 python tools/stress_det.py tiny $p 400 & done; wait
  for i in 1 2; do timeout 600 python tools/stress_det.py eurlex4k $p 300 & done; wait
done 2>&1 | grep -v Warning
