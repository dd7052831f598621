python paper_conf_cgo_shobakimhlmkrg24_b200/build.py > /dev/null
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -4
AB_ENVS="ACO_LEAN=0 ACO_LEAN=1" bash tools/ab_env.sh
