import pytest
@pytest.fixture(autouse=True)
def _ws_check(request):
    yield
    try:
        import torch, paper_conf_sc_huangd0lc23_b200 as cz
        if not torch.cuda.is_available():
            return
        torch.cuda.synchronize()
        for k, w in list(cz._ws_cache.items()):
            c = w.buf[:32].cpu().view(torch.int32).tolist()
            if c[7] != 0 or c[5] != 0 or c[6] != 0:
                print(f"\nWSCHECK after {request.node.nodeid}: ws{k} bytes={w.nbytes} ctrl={c}")
    except Exception as e:
        print("wscheck error", e)
