bash scripts/gpu_round.sh d13 tests
for wl in reddit proteins; do bash scripts/gpu_round.sh d13 bench $wl --steps 20 --warmup 5; done
bash scripts/profile_round.sh d13 reddit
for P in 2 4 8; do bash scripts/gpu_round.sh d13 solo reddit $P; done
for P in 2 4 8; do bash scripts/gpu_round.sh d13 solo proteins $P; done
