for v in new old new old; do if [ $v = old ]; then python tmp_ab/tools/gemm_ab.py old; else python tools/gemm_ab.py new; fi; done
