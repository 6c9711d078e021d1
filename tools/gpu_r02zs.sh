timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "error or large_batch or payload or append or online or snapshot or device or mixed or gids or sharded" 2>&1 | tail -3
PROBE_LIB=build/variants/at/libffm.so timeout 300 python tools/probe_append.py 2>&1 | grep "^\[append\]" | tail -7
bash tools/ab_online.sh
