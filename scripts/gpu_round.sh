set -x
CFG=c3 TAG=r01b timeout 1500 bash scripts/profile.sh
