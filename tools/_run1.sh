bash tools/profile_round.sh r01
