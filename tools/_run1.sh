timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
bash tools/profile_round.sh r01
bash tools/evidence.sh 2>&1
