bash tools/ab.sh "base:libspinfer_base.so:" "base2:libspinfer_base2.so:" "rag:libspinfer_rag.so:" "rag2:libspinfer_rag2.so:"
