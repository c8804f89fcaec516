set -x
bash tools/ncu_profile.sh r01b "prefix tuple2"
