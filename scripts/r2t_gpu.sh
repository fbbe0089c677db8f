cd $GRAFT_REPO_ROOT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "default or tm_nt1024 or tm_split or tm_static" 2>&1 | tail -2
bash scripts/ab_gpu.sh r2t "c2 c5 c3 c1" "X=0" 2
