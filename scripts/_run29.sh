bash scripts/gpu_round.sh d29 tests
for wl in reddit proteins products cora; do bash scripts/gpu_round.sh d29 bench $wl --steps 20 --warmup 5; done
for P in 2 4 8; do bash scripts/gpu_round.sh d29 solo reddit $P; done
for P in 2 4 8; do bash scripts/gpu_round.sh d29 solo proteins $P; done
