tools/ab_run.sh "rmat24 rmat24_llp" 5 base17
GLP_L2_WINDOW=1 tools/ab_run.sh "rmat24 rmat24_llp" 5 base17
python -c "
import torch; p=torch.cuda.get_device_properties(0); print('persistingL2CacheMaxSize', p.persisting_l2_cache_max_size if hasattr(p,'persisting_l2_cache_max_size') else '?', 'L2', p.L2_cache_size)"
