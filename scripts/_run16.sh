bash scripts/gpu_round.sh d16 sanitize
bash scripts/gpu_round.sh d16 tests
for P in 4; do bash scripts/gpu_round.sh d16 solo proteins $P; bash scripts/gpu_round.sh d16 solo reddit $P; done
