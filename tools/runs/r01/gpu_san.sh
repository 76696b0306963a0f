set -x
bash tools/sanitize.sh
