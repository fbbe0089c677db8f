cd $GRAFT_REPO_ROOT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "default" 2>&1 | tail -1
bash scripts/ab_gpu.sh r2v "c2 c5 c1" "SYNERGY_TM_L1PF=0 SYNERGY_TM_L1PF=1" 2
