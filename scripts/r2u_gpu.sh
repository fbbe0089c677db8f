cd $GRAFT_REPO_ROOT
python -c "from paper_conf_sc_fandccfc23_b200 import build; build.build(); import tools; tools.build()" > /dev/null 2>&1
bash scripts/ab_gpu.sh r2u "c2 c3 c4" "SYNERGY_TM_CTAS=0 SYNERGY_TM_CTAS=296 SYNERGY_TM_CTAS=444" 1
